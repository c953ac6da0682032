#!/bin/bash
# GPU tests (optionally filtered) + one C2 bench line.  Usage: bash tools/gpu_quick.sh <tag> [pytest -k expr]
TAG=${1:-quick}; OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x -p no:randomly ${2:+-k "$2"} > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
tail -3 $OUT/pytest.log
timeout 300 python bench.py --steps 10 --no-e2e --no-cpu > $OUT/bench.json 2> $OUT/bench.err
python -c "import json; d=json.load(open('$OUT/bench.json')); print(round(d['ms_per_step'],3), 'ms/step', round(d['ms_solve_per_step'],3), 'solve', round(d['roofline']['frac'],4))"
