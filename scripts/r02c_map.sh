#!/bin/bash
set -u
tag=${1:-r02cp}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_round2.py tests/test_gpu_round2c.py -q -x -k "c1_vs or medium or perm or post_modes or residue or sparse or cluster_centroid or shard or gen" > gpurun_out/${tag}_pytest.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest.txt
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -k "c5 or c2_every" >> gpurun_out/${tag}_pytest.txt 2>&1
echo "pytest2 rc=$?" >> gpurun_out/${tag}_pytest.txt
timeout 300 python bench.py --config C5 --no-cpu-baseline > gpurun_out/${tag}_C5.json 2> gpurun_out/${tag}_C5.err
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-general > gpurun_out/${tag}_C2.json 2> gpurun_out/${tag}_C2.err
P="python scripts/profile_step.py"
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${tag}_launches_C2t10.csv $P --config C2 --t 10 > /dev/null 2>&1
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_res "map_dist|residual_traj" 0 2 $P --config C2 --t 10
ls gpurun_out | grep $tag
