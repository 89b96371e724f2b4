# One gpurun call: GPU tests, the default bench line, the reference arm, the
# ncu launch list of the timed configuration only (--profile: no e2e, no CPU
# baseline, no parity tail), and one ncu --set full capture of the bench's
# replay kernel (compact lane-per-trace, one launch per policy).
# Usage: bash scripts/profile_round.sh <tag>
set -x
T=${1:-r02}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python bench.py --steps 3 --warmup 3 --profile > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu_launch=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_lpt16 -c 4 -o gpurun_out/${T}_prof python bench.py --steps 1 --warmup 1 --profile > gpurun_out/ncu_full.log 2>&1; echo ncu_full=$?
ls -la gpurun_out
