# Tuning call for the NEXT-3 wrapper kernel: its parity tests on the current
# build, then the wrap bench (HBM GB/s) of ab/base.so and ab/wrap_new.so.
timeout 900 python -m pytest tests/test_gpu_wrap.py -x -q > gpurun_out/pytest_wrap.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_wrap.log
for r in 1 2; do for so in base wrap_new; do
  CONVGPU_SO=ab/$so.so timeout 300 python scripts/wrap_bench.py 2>/dev/null | tail -1 > gpurun_out/wrap_$so.json
  python -c "import json; d=json.load(open('gpurun_out/wrap_$so.json')); r=d.get('roofline', d); print('$so', {k: r[k] for k in r if k in ('achieved','frac','unit')} , d.get('value'))"
done; done
