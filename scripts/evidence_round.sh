# Round-end evidence in one gpurun call: GPU tests, smoke, the default bench
# line, the reference arm, config [1] / paper-mimic / config [3] lines, the
# launch list of the timed configuration and one ncu --set full capture of
# the bench's replay kernel.   Usage: bash scripts/evidence_round.sh <tag>
set -x
T=${1:-r02}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
if [ -z "$SKIP_PYTEST" ]; then timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${T}_pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/${T}_pytest_gpu.log; fi
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo smoke=$?
timeout 600 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo bench=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${T}_bench_ref.json 2> gpurun_out/${T}_bench_ref.err; echo ref=$?
timeout 600 python bench.py --workload c1 --no-cpu-baseline > gpurun_out/${T}_bench_c1.json 2> gpurun_out/${T}_bench_c1.err; echo c1=$?
timeout 600 python bench.py --workload mimic --no-cpu-baseline > gpurun_out/${T}_bench_mimic.json 2> gpurun_out/${T}_bench_mimic.err; echo mimic=$?
timeout 900 python bench.py --workload c3 --steps 2 --warmup 1 > gpurun_out/${T}_bench_c3.json 2> gpurun_out/${T}_bench_c3.err; echo c3=$?
timeout 900 python scripts/rho_sweep.py --out gpurun_out/${T}_rho_sweep.json > gpurun_out/${T}_rho_sweep.txt 2>&1; echo rho=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python bench.py --steps 3 --warmup 3 --profile > gpurun_out/ncu_launch_bench.log 2>&1; echo ncu_launch=$?
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:replay_lpt16_kernel<.*bool.0>' -c 4 -o gpurun_out/${T}_prof python bench.py --steps 1 --warmup 1 --profile > gpurun_out/ncu_full.log 2>&1; echo ncu_full=$?
# summarise on the box (the report itself can exceed gpurun's 64 MiB copy-back)
mkdir -p gpurun_out/summ
NCU_SUMMARY_DIR=gpurun_out/summ python scripts/summarize_ncu.py --rep gpurun_out/${T}_prof.ncu-rep --tag ${T} --traffic --only 'replay_lpt16_kernel<\(int\)\d, \(bool\)0>|replay_lpt16_kernel<\d, 0>' > gpurun_out/summ.log 2>&1; echo summ=$?
ncu -i gpurun_out/${T}_prof.ncu-rep --page source --csv --print-source sass > /tmp/${T}_src.csv 2>/dev/null; gzip -c /tmp/${T}_src.csv > gpurun_out/${T}_src.csv.gz
mv gpurun_out/${T}_prof.ncu-rep /tmp/ 2>/dev/null
ls -la gpurun_out
