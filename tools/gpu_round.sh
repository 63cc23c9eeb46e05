#!/bin/bash
# One GPU session: parity tests, full sweep, bench, ncu launch list + full captures.
# Usage (under gpurun): bash tools/gpu_round.sh <tag>
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi_$TAG.txt
timeout 900 python -m pytest tests -m gpu -q -rf --timeout 900 > $O/pytest_gpu_$TAG.log 2>&1; echo PYTEST_RC=$? >> $O/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo SMOKE_RC=$? >> $O/smoke_$TAG.log
timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err
timeout 600 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo BENCH_RC=$? >> $O/bench_$TAG.err
timeout 120 python tools/resource_table.py $TAG > /dev/null 2>&1
timeout 1500 python tools/sweep.py --out $O/sweep_$TAG.jsonl > $O/sweep_$TAG.log 2>&1; echo SWEEP_RC=$? >> $O/sweep_$TAG.log
TCFG=$(python -c "import json;d=json.load(open('$O/bench_$TAG.json'));c=d['config']['tmv'];print(f\"{c['S']},{c['dist']},{c['map']}\")" 2>/dev/null || echo 32,block,inter)
MCFG=$(python -c "import json;d=json.load(open('$O/bench_$TAG.json'));c=d['config']['mv'];print(f\"{c['S']},{c['dist']},{c['map']}\")" 2>/dev/null || echo 32,cyclic,intra)
echo "TCFG=$TCFG MCFG=$MCFG" > $O/cfg_$TAG.txt
# the launch list of the driver's own command (default `python bench.py`), and of the timed
# step alone (--no-sweep: the two kernels of the step and the input generator)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_full_$TAG.csv python bench.py > $O/bench_ncu_full_$TAG.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv python bench.py --steps 5 --warmup 2 --no-cpu-baseline --e2e-steps 0 --no-sweep --tmv-cfg $TCFG --mv-cfg $MCFG > $O/bench_ncu_$TAG.log 2>&1
IFS=, read TS TD TM <<< "$TCFG"
IFS=, read MS MD MM <<< "$MCFG"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tmv_ -s 2 -c 1 -o $O/prof_tmv_$TAG python tools/ncu_target.py --op tmv --S $TS --dist $TD --map $TM > $O/ncu_tmv_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:mv_ -s 2 -c 1 -o $O/prof_mv_$TAG python tools/ncu_target.py --op mv --S $MS --dist $MD --map $MM > $O/ncu_mv_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:reduce_ -s 2 -c 1 -o $O/prof_reduce_$TAG python tools/ncu_target.py --op reduce --S 8 --dist block --map intra --L 64 > $O/ncu_reduce_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:scan_ -s 2 -c 1 -o $O/prof_scan_$TAG python tools/ncu_target.py --op scan --S 16 --dist cyclic --map intra --L 256 --N 2097152 --dtype i32 > $O/ncu_scan_$TAG.log 2>&1
ls $O
