# Tuning call: A/B times of ab/*.so on config [2], plus one ncu --set full
# capture of the FIFO and Best-Fit compact-kernel launches (pipe utilisation,
# instruction mix) of the current build.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
bash scripts/ab_time.sh 2>&1 | tee gpurun_out/ab.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:replay_lpt16 -c 2 -o gpurun_out/probe python scripts/exp_lpt.py --kernel lane16 --env X --values 0 --reps 1 > gpurun_out/probe.log 2>&1; echo ncu=$?
