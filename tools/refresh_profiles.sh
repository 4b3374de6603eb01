# Run on the GPU box (gpurun): the default bench line, the ncu launch list of the same command, and one
# --set full capture of each hot kernel. Outputs land in gpurun_out/; summarise them into profiles/
# here with tools/ncu_summary.py (see profiles/README in DESIGN.md §8).
set -x
python bench.py > gpurun_out/bench_line.log 2> gpurun_out/bench_err.log
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-configs > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:'k_search_r1|k_eval|k_switch|k_search_generic' -c 8 \
  -o gpurun_out/kernels_full python tools/profile_kernels.py > gpurun_out/profile_kernels.log 2>&1
ls -la gpurun_out
