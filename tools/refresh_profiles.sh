# Run on the GPU box (gpurun): the default bench line, the ncu launch list of the same command, one
# --set full capture of each hot kernel (summarised on the box; the report itself is too large to
# bring back), the per-kernel DRAM traffic, and a source-annotated capture of the hot search kernel.
# Outputs land in gpurun_out/; copy the summaries into profiles/ here (round-named).
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python bench.py > gpurun_out/bench_line.log 2> gpurun_out/bench_err.log
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-configs --secondary '' > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/launches.csv > gpurun_out/launches_summary.txt
ncu --set full --clock-control none -k regex:'k_search_r1|k_eval|k_switch|k_search_dfs|k_search_generic|k_search_rr|k_rr_drain' -c 48 \
  -o /tmp/kernels_full python tools/profile_kernels.py > gpurun_out/profile_kernels.log 2>&1
python tools/ncu_summary.py full /tmp/kernels_full.ncu-rep > gpurun_out/kernels_full.txt
python tools/ncu_summary.py traffic /tmp/kernels_full.ncu-rep > gpurun_out/traffic.json
ls -la gpurun_out
