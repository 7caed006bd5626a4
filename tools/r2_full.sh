#!/bin/bash
# full GPU check: all GPU tests, the bench line, the ladder ncu captures
mkdir -p gpurun_out/full
export PYTHONUNBUFFERED=1
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/full/pytest.txt 2>&1; tail -4 gpurun_out/full/pytest.txt
timeout 1200 python bench.py > gpurun_out/full/bench.json 2> gpurun_out/full/bench.err; echo "bench rc=$?"; tail -3 gpurun_out/full/bench.err
[ -n "$LADDER" ] && bash tools/ladder_ncu.sh
