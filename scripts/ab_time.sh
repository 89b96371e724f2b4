# Time every ab/*.so on config [2] (lane16), interleaved, two rounds.
for r in 1 2; do for f in ab/*.so; do
  echo -n "$(basename $f .so) "; CONVGPU_SO=$f timeout 200 python scripts/exp_lpt.py --kernel ${KERNEL:-lane16} --env X --values 0 2>&1 | tail -1
done; done
