# Kernel time of the full 96-layer search (both states) and of one 8-way shard, per library variant
# (LIBS = in-tree .so names built with different compile-time options).
for lib in ${LIBS:-libautopipe.so}; do
  for kind in a-nvlink b; do
    echo "$lib $(AUTOPIPE_LIB=$PWD/paper_conf_icpp_hulww24_b200/$lib python tools/one_shard.py $kind 1 0) | $(AUTOPIPE_LIB=$PWD/paper_conf_icpp_hulww24_b200/$lib python tools/one_shard.py $kind 8 7)"
  done
done
