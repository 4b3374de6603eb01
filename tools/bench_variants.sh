for lib in ${LIBS:-libautopipe.so}; do
  AUTOPIPE_LIB=$PWD/paper_conf_icpp_hulww24_b200/$lib timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', round(d['ms_per_step'],3), round(d['value']/1e9,1), d['secondary_states']['b']['ms_per_step'], d['optimum'], d['secondary_states']['b']['optimum_T_ns'])"
done
