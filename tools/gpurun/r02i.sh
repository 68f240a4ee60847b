timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -4
timeout 300 python tools/quick_time.py C2 2>&1 | grep -E "SSIM|ALL"
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1500 compute-sanitizer --tool initcheck --print-limit 50 python tools/sanitize_target.py > gpurun_out/sanitize_initcheck_r02.log 2>&1; tail -2 gpurun_out/sanitize_initcheck_r02.log
