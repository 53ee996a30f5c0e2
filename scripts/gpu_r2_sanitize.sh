# compute-sanitizer memcheck / racecheck / synccheck of the library's kernels (profiles/r02_sanitizer_*.log)
python -c "import __graft_entry__ as g; g.build()" || exit 1
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck --leak-check full --print-limit 50 python scripts/sanitize_driver.py all > gpurun_out/r02_sanitizer_memcheck.log 2>&1; echo "memcheck rc=$?"
timeout 1500 $CS --tool racecheck --print-limit 50 python scripts/sanitize_driver.py tiny > gpurun_out/r02_sanitizer_racecheck.log 2>&1; echo "racecheck rc=$?"
timeout 1500 $CS --tool synccheck --print-limit 50 python scripts/sanitize_driver.py tiny > gpurun_out/r02_sanitizer_synccheck.log 2>&1; echo "synccheck rc=$?"
tail -3 gpurun_out/r02_sanitizer_*.log
