timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "lane" 2>&1 | tail -2
for k in lane warp; do timeout 300 python bench.py --kernel $k --steps 3 --warmup 1 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['kernel'], '%.3g'%d['value'], {p:round(v['launch_ms'],2) for p,v in d['per_policy'].items()})"; done
