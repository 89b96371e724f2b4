set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:replay_lpt16 -c 4 -o gpurun_out/prof_r02a python bench.py --steps 1 --warmup 1 --profile --no-check > gpurun_out/ncu_full.log 2>&1; echo ncu=$?
ls -la gpurun_out
