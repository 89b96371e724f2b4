# Tuning call for the NEXT-3 wrapper kernel: its parity tests on the current
# build, then the wrap bench (HBM GB/s) of every ab/*.so.
timeout 900 python -m pytest tests/test_gpu_wrap.py -x -q > gpurun_out/pytest_wrap.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_wrap.log
for r in 1 2; do for f in ab/*.so; do so=$(basename $f .so)
  CONVGPU_SO=$f timeout 300 python scripts/wrap_bench.py 2>/dev/null | tail -1 > gpurun_out/wrap_$so.json
  python -c "import json; d=json.load(open('gpurun_out/wrap_$so.json')); r=d.get('roofline', d); print('$so', round(r['achieved']), round(r['frac'], 3))"
done; done
