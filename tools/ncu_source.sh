# Source-level ncu capture of one kernel of tools/profile_one.py (run on the GPU box via gpurun):
#   bash tools/ncu_source.sh <workload> <kernel-regex> <name>
# writes gpurun_out/<name>.ncu-rep, <name>_sass.csv and <name>_summary.txt
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"$2" -c 1 -o gpurun_out/$3 \
  python tools/profile_one.py $1 > gpurun_out/$3_run.log 2>&1
ncu -i gpurun_out/$3.ncu-rep --page source --csv --print-source sass > gpurun_out/$3_sass.csv 2>&1
python tools/ncu_summary.py full gpurun_out/$3.ncu-rep > gpurun_out/$3_summary.txt 2>&1
