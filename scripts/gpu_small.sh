# AUTO threshold data: per-policy launch time of each replay kernel at small
# batch sizes (config [2] traces).
for n in 1000 2000 4736 9472 16960; do for k in warp lane lane16; do
  echo -n "n=$n "; timeout 200 python scripts/exp_lpt.py --kernel $k --env X --values 0 --traces $n 2>&1 | tail -1
done; done
