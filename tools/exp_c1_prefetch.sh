#!/bin/bash
# A/B of the narrow TMV's L2 prefetch before griddepcontrol.wait on C1 (graph of
# 64 cold launches): default library vs a -DCUDANP_TMV_PREFETCH=0 build.
# Usage (under gpurun): bash tools/exp_c1_prefetch.sh <tag>
TAG=${1:-c1pf}
O=gpurun_out
mkdir -p $O
NOPF=paper_conf_ppopp_yangz14_b200/libcudanp_nopf.so
[ -f $NOPF ] || python -m paper_conf_ppopp_yangz14_b200.build -DCUDANP_TMV_PREFETCH=0 --out $NOPF
for rep in 1 2; do
  echo "{\"variant\": \"prefetch\", \"rep\": $rep, \"r\": $(python tools/exp_c1_warm.py)}" >> $O/exp_c1pf_$TAG.jsonl
  echo "{\"variant\": \"no_prefetch\", \"rep\": $rep, \"r\": $(CUDANP_LIB=$NOPF python tools/exp_c1_warm.py)}" >> $O/exp_c1pf_$TAG.jsonl
done
python tools/c1_latency.py --out $O/c1_latency_$TAG.jsonl > /dev/null 2>&1
cat $O/exp_c1pf_$TAG.jsonl
