#!/bin/bash
# Round-2 ncu captures (GPU box, repo root); outputs gpurun_out/<tag>_*:
#   launch list of one C3 step; --set full of the C3 row-resident kernel; --set full of map_residual and
#   the residue trajectory kernel at C2 t=10; --set full of one general-CSC (ELL) layer launch at C2 perm.
set -u
tag=$1
mkdir -p gpurun_out
P="python scripts/profile_step.py"
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C3.csv $P --config C3 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_C3 pre_fused 0 1 $P --config C3
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_res "map_residual|residual_traj" 0 2 $P --config C2 --t 10
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C2t10.csv $P --config C2 --t 10 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_ell layer_ell 2 1 $P --config C2 --mode perm
ls -la gpurun_out/ | grep $tag
