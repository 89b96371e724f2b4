nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python scripts/exp_skip_check.py --ref ab_ref/head.so --var ab/base.so > gpurun_out/check_base.txt 2>&1; echo check_base=$?; tail -4 gpurun_out/check_base.txt
timeout 300 python scripts/exp_skip_check.py --ref ab_ref/head.so --var ab/skip.so --ignore peak_used,digest > gpurun_out/check_skip.txt 2>&1; echo check_skip=$?; tail -4 gpurun_out/check_skip.txt
cp ab_ref/head.so ab/head.so
bash scripts/ab_time.sh 2>&1 | tee gpurun_out/ab.txt
