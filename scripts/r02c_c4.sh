#!/bin/bash
# Round 2 (r02c): general-CSC kernel + cluster R30 check (GPU box, repo root).  Outputs gpurun_out/<tag>_*.
set -u
tag=${1:-r02cj}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_round2c.py tests/test_gpu_parity.py tests/test_gpu_round2.py -q -x -k "gen or ell or perm or medium or ragged or random or uncompressed or post_modes or pre_fused or range or cluster" > gpurun_out/${tag}_pytest.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/${tag}_pytest.txt
timeout 300 python bench.py --config C2 --mode perm --quick --no-cpu-baseline > gpurun_out/${tag}_C2perm.json 2> gpurun_out/${tag}_C2perm.err
timeout 300 python bench.py --config C5 --t 18 --quick --no-cpu-baseline > gpurun_out/${tag}_C5u.json 2> gpurun_out/${tag}_C5u.err
timeout 300 python bench.py --config C5 --quick --no-cpu-baseline > gpurun_out/${tag}_C5.json 2> gpurun_out/${tag}_C5.err
timeout 400 python bench.py --config C4 --quick --no-cpu-baseline --pre-fused 4 > gpurun_out/${tag}_C4pf4.json 2> gpurun_out/${tag}_C4pf4.err
timeout 400 python bench.py --config C4 --quick --no-cpu-baseline > gpurun_out/${tag}_C4.json 2> gpurun_out/${tag}_C4.err
timeout 300 python bench.py --config C3 --quick --no-cpu-baseline --pre-fused 4 > gpurun_out/${tag}_C3pf4.json 2> gpurun_out/${tag}_C3pf4.err
NCU_EXTRA="--profile-from-start off" scripts/ncu_capture.sh ${tag}_full_gen5 layer_gen 2 1 python scripts/profile_step.py --config C5 --t 18
ls gpurun_out | grep $tag
