#!/bin/bash
# Round measurement suite for one config (run on the GPU box from the repo root):
#   scripts/measure.sh <tag> <config> [bench args...]
# -> gpurun_out/<tag>_bench.json      bench.py line (default flags + extra args)
#    gpurun_out/<tag>_launches.csv    ncu launch list of one step (gpu__time_duration, clock-control none)
#    gpurun_out/<tag>_traffic.csv     ncu dram read/write bytes of the a1 kernels of one step
#    gpurun_out/<tag>_full.*.csv      ncu --set full of the first a1 launch(es)
# PF=0 profiles the per-layer kernels (layer_circ*), else the row-resident pre_fused_kernel.
set -u
tag=$1; cfg=$2; shift 2
PF=${PF:-1}
if [ "$PF" = "0" ]; then kre="layer_circ"; nfull=3; else kre="pre_fused"; nfull=1; fi
mkdir -p gpurun_out
python bench.py --config "$cfg" --pre-fused "$PF" "$@" > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches.csv python scripts/profile_step.py --config "$cfg" --pre-fused "$PF" > /dev/null 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    --profile-from-start off -k regex:$kre --csv --log-file gpurun_out/${tag}_traffic.csv \
    python scripts/profile_step.py --config "$cfg" --pre-fused "$PF" > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full "$kre" 0 $nfull \
    python scripts/profile_step.py --config "$cfg" --pre-fused "$PF"
