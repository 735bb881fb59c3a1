#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
run() { # name, case, hints
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 -o gpurun_out/$1 python tools/sweep.py --case $2 --reps 1 --hints "$3" > gpurun_out/$1.log 2>&1
}
run p_od32x128 5120,5120:1,0:8 '{"schema":"OD","in_dim":0,"in_block":32,"out_dim":0,"out_block":128}'
run p_od64x64 5120,5120:1,0:8 '{"schema":"OD","in_dim":0,"in_block":64,"out_dim":0,"out_block":64}'
run p_oa2049 16,20,16,20,16,16:2,0,4,1,5,3:8 '{"schema":"OA","in_dim":1,"in_block":20,"out_dim":1,"out_block":16}'
run p_od2007 320,320,256:1,0,2:8 '{"schema":"OD","in_dim":0,"in_block":16,"out_dim":0,"out_block":320}'
python tools/sweep.py --case 5120,5120:1,0:8 --reps 10 --hints '{"schema":"OD","in_dim":0,"in_block":32,"out_dim":0,"out_block":128}' --hints '{"schema":"OD","in_dim":0,"in_block":32,"out_dim":0,"out_block":128,"variant":2}' --hints '{"schema":"OD","in_dim":0,"in_block":64,"out_dim":0,"out_block":64}' --hints '{"schema":"OD","in_dim":0,"in_block":64,"out_dim":0,"out_block":64,"variant":2}' --hints '{"schema":"OD","in_dim":0,"in_block":32,"out_dim":0,"out_block":256,"variant":1}' --hints '{"schema":"OD","in_dim":0,"in_block":64,"out_dim":0,"out_block":128,"variant":1}' --hints '{"schema":"OD","in_dim":0,"in_block":128,"out_dim":0,"out_block":64,"variant":1}' --hints '{"schema":"OD","in_dim":0,"in_block":16,"out_dim":0,"out_block":256}' --hints '{"schema":"OD","in_dim":0,"in_block":256,"out_dim":0,"out_block":16}' > gpurun_out/sweep3.jsonl 2>&1
