timeout 900 python -m pytest tests/test_gpu_lane16.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_sp.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_sp.log
for r in 1 2; do for so in base spread; do
  CONVGPU_SO=ab/$so.so timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 5 2>/dev/null | tail -1 > gpurun_out/sp_$so.json
  python -c "import json; d=json.load(open('gpurun_out/sp_$so.json')); print('$so value %.3e e2e %.3e' % (d['value'], d['e2e']['value']))"
done; done
for so in base spread; do CONVGPU_SO=ab/$so.so timeout 200 python scripts/exp_lpt.py --kernel lane16 --env X --values 0 --traces 32768 2>&1 | tail -1; CONVGPU_SO=ab/$so.so timeout 200 python scripts/exp_lpt.py --kernel lane16 --env X --values 0 --traces 20000 2>&1 | tail -1; done
