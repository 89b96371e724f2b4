# One gpurun call while tuning the compact kernel: its parity tests, then the
# per-policy launch times on config [2].
timeout 700 python -m pytest tests/test_gpu_lane16.py -x -q > gpurun_out/pytest_lane16.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_lane16.log
timeout 200 python scripts/exp_lpt.py --kernel lane16 --env X --values 0 2>&1 | tail -2
