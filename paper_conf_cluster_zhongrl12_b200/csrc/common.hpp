// Shared error plumbing of libfpmpmm (no CUDA types here).
#pragma once

#include <cstdarg>
#include <cstdint>
#include <exception>
#include <string>

#include "fpmpmm.h"

namespace fpm {

// Thrown inside the library, converted to a status code at the ABI boundary.
struct Error : std::exception {
    int code;
    std::string msg;
    Error(int c, std::string m) : code(c), msg(std::move(m)) {}
    const char* what() const noexcept override { return msg.c_str(); }
};

void set_last_error(const std::string& msg);
[[noreturn]] void fail(int code, const char* fmt, ...) __attribute__((format(printf, 2, 3)));

#define FPM_CHECK_ARG(cond, ...)                          \
    do {                                                  \
        if (!(cond)) ::fpm::fail(FPM_EINVAL, __VA_ARGS__); \
    } while (0)

// Run `body` and translate exceptions into status codes (the ABI boundary).
template <class F>
int guarded(F&& body) {
    try {
        body();
        return FPM_OK;
    } catch (const Error& e) {
        set_last_error(e.msg);
        return e.code;
    } catch (const std::bad_alloc&) {
        set_last_error("host allocation failed");
        return FPM_ENOMEM;
    } catch (const std::exception& e) {
        set_last_error(std::string("internal error: ") + e.what());
        return FPM_EINVAL;
    }
}

}  // namespace fpm
