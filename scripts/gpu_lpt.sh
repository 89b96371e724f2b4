set -x
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -15 gpurun_out/pytest_gpu.log
for k in lane warp; do timeout 300 python bench.py --kernel $k --steps 10 --no-e2e --no-cpu-baseline > gpurun_out/bench_$k.json 2> gpurun_out/bench_$k.err; echo bench_$k=$?; tail -2 gpurun_out/bench_$k.err; done
