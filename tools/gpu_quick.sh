#!/bin/bash
# Quick GPU check: parity tests + sweep of the given configs (+ optional bench).
# Usage (under gpurun): bash tools/gpu_quick.sh <tag> <configs> [bench]
TAG=${1:-q}; CFGS=${2:-C2}; O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -rf --timeout 900 > $O/pytest_gpu_$TAG.log 2>&1; echo PYTEST_RC=$? >> $O/pytest_gpu_$TAG.log
timeout 900 python tools/sweep.py --configs $CFGS --out $O/sweep_$TAG.jsonl > $O/sweep_$TAG.log 2>&1
if [ "$3" = "bench" ]; then timeout 600 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; fi
tail -2 $O/pytest_gpu_$TAG.log
