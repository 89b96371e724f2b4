# One gpurun call: GPU tests, the default bench line, the reference arm, the
# ncu launch list of the bench command, and one ncu --set full capture of the
# bench's replay kernel (compact lane-per-trace, one launch per policy).
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu_launch=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_lpt16 -c 4 -o gpurun_out/prof_lane16 python bench.py --steps 1 --warmup 1 --profile > gpurun_out/ncu_full_lane16.log 2>&1; echo ncu_lane16=$?
ls -la gpurun_out
