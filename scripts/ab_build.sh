# Build the current csrc/ into ab/<name>.so for an A/B timing run
# (scripts/ab_time.sh); ab/ travels with the gpurun snapshot (*.so is git-ignored).
set -e
cd "$(dirname "$0")/.."
python -c "from paper_conf_cluster_kangjkkk17_b200 import build as b; b.build(force=True)" >/dev/null
cp paper_conf_cluster_kangjkkk17_b200/libconvgpu.so ab/$1.so
