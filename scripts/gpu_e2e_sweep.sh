# Tuning call: the end-to-end (host-buffer) rate of bench.py over chunk sizes,
# interleaved repetitions (the host path is copy-bound and noisy).
for r in 1 2 3; do for c in 32768 65536 131072; do
  timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 5 --e2e-chunk $c 2>/dev/null | tail -1 > gpurun_out/e2e_$c.json
  python -c "import json,sys; d=json.load(open('gpurun_out/e2e_$c.json')); print('chunk $c', 'value %.3e' % d['value'], 'e2e %.3e' % d['e2e']['value'])"
done; done
