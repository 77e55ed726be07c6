#!/bin/bash
# round-2 batch 3: the paired coarse-group sorts of the B-Limited kernel -- parity (limited paths,
# whole C3 / C5) and the C2 / C3 / C5 lines
cd $GRAFT_REPO_ROOT
python -m pytest tests/test_gpu_parity.py -x -q -k "limited or zeros or overflow or c_matches or tiny or clustered" 2>&1 | tail -2 > gpurun_out/b3_pytest.txt
python -m pytest tests/test_gpu_full.py -x -q -k "C3-opts3 or C5-opts5" 2>&1 | tail -2 >> gpurun_out/b3_pytest.txt
python bench.py --config C2 --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/b_c2.json 2>&1
python bench.py --config C3 --no-e2e --no-cpu-baseline --steps 3 > gpurun_out/b_c3.json 2>&1
python bench.py --config C5 --no-e2e --no-cpu-baseline --steps 3 > gpurun_out/b_c5.json 2>&1
cat gpurun_out/b3_pytest.txt
