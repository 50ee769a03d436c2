# Build an experiment variant of libffs.so into exp/<name>.so (git-ignored; travels with gpurun).
#   bash tools/build_variant.sh <name> [nvcc -D flags ...]
set -e
cd "$(dirname "$0")/.."
name=$1; shift
C=paper_conf_hpdc_hui0s25_b200/csrc
mkdir -p exp
/usr/local/cuda/bin/nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC -shared \
  -Iinclude "$@" -o exp/$name.so $C/ffs_host.cu $C/ffs_kernels.cu
