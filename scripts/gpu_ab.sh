# Tuning call: parity of the current build (compact-kernel tests), then A/B
# times of every ab/*.so on config [2].
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 700 python -m pytest tests/test_gpu_lane16.py -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_lane16.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_lane16.log
bash scripts/ab_time.sh 2>&1 | tee gpurun_out/ab.txt
