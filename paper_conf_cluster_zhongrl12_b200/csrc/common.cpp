#include "common.hpp"

#include <cstdio>

namespace fpm {

static thread_local std::string g_last_error = "no error";

void set_last_error(const std::string& msg) { g_last_error = msg; }

void fail(int code, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    std::vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    throw Error(code, buf);
}

}  // namespace fpm

extern "C" const char* fpm_last_error(void) { return fpm::g_last_error.c_str(); }
extern "C" int32_t fpm_abi_version(void) { return 1; }
