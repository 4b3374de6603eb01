# Build in-tree variants of libautopipe.so with different compile-time options of the hot kernel
# (for tools/variant_times.sh): each argument is NAME=FLAGS, e.g. "v4nx2=-DR1_V4=1 -DR1_NX=2".
set -e
cd "$(dirname "$0")/../paper_conf_icpp_hulww24_b200/csrc"
for spec in "$@"; do
  name="${spec%%=*}"; flags="${spec#*=}"
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared $flags \
    -o ../libautopipe_${name}.so autopipe.cu kernels.cu &
done
wait
