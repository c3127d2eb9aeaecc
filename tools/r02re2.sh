O=gpurun_out/r02re2; mkdir -p $O
timeout 300 python tools/sanitize_r02b.py > $O/plain.log 2>&1; echo "rc=$?" >> $O/plain.log
timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_r02b.py > $O/san_memcheck.log 2>&1; echo "rc=$?" >> $O/san_memcheck.log
timeout 1200 compute-sanitizer --tool racecheck python tools/sanitize_r02b.py > $O/san_racecheck.log 2>&1; echo "rc=$?" >> $O/san_racecheck.log
timeout 1200 compute-sanitizer --tool synccheck python tools/sanitize_r02b.py > $O/san_synccheck.log 2>&1; echo "rc=$?" >> $O/san_synccheck.log
