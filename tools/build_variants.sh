# Build in-tree variants of libautopipe.so with different compile-time options (for timing
# experiments; select one with AUTOPIPE_LIB=<path>): each argument is NAME=FLAGS, e.g.
# "per8=-DEVAL_PER16=8". TUS (default: all) names the translation units compiled with the flags;
# the others are linked from the regular build (paper_conf_icpp_hulww24_b200/build/*.o).
set -e
cd "$(dirname "$0")/../paper_conf_icpp_hulww24_b200/csrc"
mkdir -p ../build/variants
ALL="autopipe k_state k_eval k_search k_search_r1 k_neigh k_switch"
TUS="${TUS:-$ALL}"
for spec in "$@"; do
  name="${spec%%=*}"; flags="${spec#*=}"
  (
    objs=""
    for f in $ALL; do
      if [[ " $TUS " == *" $f "* ]]; then
        nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC $flags \
          -c -o ../build/variants/${name}_$f.o $f.cu &
        objs="$objs ../build/variants/${name}_$f.o"
      else
        objs="$objs ../build/$f.o"
      fi
    done
    wait
    nvcc -gencode arch=compute_100a,code=sm_100a -shared -o ../libautopipe_${name}.so $objs
  ) &
done
wait
