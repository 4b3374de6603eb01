# Run on the GPU box (gpurun): the default bench line, the ncu launch list of the same command, one
# --set full capture of each hot kernel (summarised on the box; the report itself is too large to
# bring back) and a source-annotated capture of the hot search kernel alone (k_search_r1<8, u32>).
# Outputs land in gpurun_out/; copy the summaries into profiles/ here.
set -x
python bench.py > gpurun_out/bench_line.log 2> gpurun_out/bench_err.log
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-configs > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/launches.csv > gpurun_out/launches_summary.txt
ncu --set full --clock-control none -k regex:'k_search_r1|k_eval|k_switch|k_search_generic' -c 8 \
  -o /tmp/kernels_full python tools/profile_kernels.py > gpurun_out/profile_kernels.log 2>&1
python tools/ncu_summary.py full /tmp/kernels_full.ncu-rep > gpurun_out/kernels_full.txt
ncu --set full --clock-control none --import-source on -k regex:'k_search_r1' -c 1 \
  -o gpurun_out/r1_u32 python tools/profile_kernels.py > /dev/null 2>&1
ncu -i gpurun_out/r1_u32.ncu-rep --page source --csv --print-source sass > gpurun_out/r1_u32_sass.csv 2>&1
ncu -i gpurun_out/r1_u32.ncu-rep --page source --csv --print-source cuda > gpurun_out/r1_u32_cuda.csv 2>&1
du -sh gpurun_out/*
# keep the pull under gpurun's 64 MiB cap
for f in gpurun_out/*; do [ "$(du -m "$f" | cut -f1)" -gt 40 ] && rm -f "$f"; done
ls -la gpurun_out
