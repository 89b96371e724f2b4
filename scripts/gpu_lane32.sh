# Tuning call for the 32-bit lane kernel: GPU parity suite on the current
# build, then A/B times of ab/*.so on config [2] with kernel=lane.
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lane16.py -x -q > gpurun_out/pytest_l32.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_l32.log
for r in 1 2; do for f in ab/*.so; do
  echo -n "$(basename $f .so) "; CONVGPU_SO=$f timeout 200 python scripts/exp_lpt.py --kernel lane --env X --values 0 2>&1 | tail -1
done; done
