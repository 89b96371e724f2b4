# Build the current csrc/ into ab/<name>.so for an A/B timing run
# (scripts/ab_time.sh); ab/ travels with the gpurun snapshot (*.so is git-ignored).
# CONVGPU_NVCC_DEFS selects a variant; the in-tree library is rebuilt without
# them afterwards, so an experiment build never stays in place.
set -e
cd "$(dirname "$0")/.."
python -c "from paper_conf_cluster_kangjkkk17_b200 import build as b; b.build(force=True)" >/dev/null
cp paper_conf_cluster_kangjkkk17_b200/libconvgpu.so ab/$1.so
if [ -n "$CONVGPU_NVCC_DEFS" ]; then
  CONVGPU_NVCC_DEFS= python -c "from paper_conf_cluster_kangjkkk17_b200 import build as b; b.build(force=True)" >/dev/null
fi
