python -m pytest tests/test_gpu_tall.py tests/test_gpu_apps.py -q 2>&1 | tail -2
python tools/kprof_orth.py 2>&1 | grep -v Warn | head -4
