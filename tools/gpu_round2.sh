#!/bin/bash
# Round-2 GPU evidence session: parity tests, smoke, both bench arms, oracle
# timing, full sweep, ncu launch lists (the driver's command and the timed step
# with the bench's own versions pinned), full captures of the timed kernels and
# the tiled S=1 baselines, compute-sanitizer.
# Usage (under gpurun): bash tools/gpu_round2.sh <tag> [quick]
TAG=${1:-r02}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi_$TAG.txt
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 1500 --durations=20 > $O/pytest_gpu_$TAG.log 2>&1; echo PYTEST_RC=$? >> $O/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo SMOKE_RC=$? >> $O/smoke_$TAG.log
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo BENCH_RC=$? >> $O/bench_$TAG.err
TCFG=$(python -c "import json;d=json.load(open('$O/bench_$TAG.json'));c=d['config']['tmv'];print(f\"{c['S']},{c['dist']},{c['map']}\")" 2>/dev/null || echo 8,cyclic,inter_tma)
MCFG=$(python -c "import json;d=json.load(open('$O/bench_$TAG.json'));c=d['config']['mv'];print(f\"{c['S']},{c['dist']},{c['map']}\")" 2>/dev/null || echo 256,cyclic,intra)
echo "TCFG=$TCFG MCFG=$MCFG" > $O/cfg_$TAG.txt
# launch list of the timed step with the bench's own versions pinned
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 0 --no-sweep --no-c5 --tmv-cfg $TCFG --mv-cfg $MCFG > $O/bench_ncu_$TAG.log 2>&1
IFS=, read TS TD TM <<< "$TCFG"
IFS=, read MS MD MM <<< "$MCFG"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tmv_ -s 2 -c 1 -o $O/prof_tmv_$TAG python tools/ncu_target.py --op tmv --S $TS --dist $TD --map $TM > $O/ncu_tmv_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:mv_ -s 2 -c 1 -o $O/prof_mv_$TAG python tools/ncu_target.py --op mv --S $MS --dist $MD --map $MM > $O/ncu_mv_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:mv_s1 -s 2 -c 1 -o $O/prof_mvtiled_$TAG python tools/ncu_target.py --op mv_tiled > $O/ncu_mvtiled_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:scan_s1 -s 2 -c 1 -o $O/prof_scantiled_$TAG python tools/ncu_target.py --op scan_tiled --L 256 --N 2097152 --dtype i32 > $O/ncu_scantiled_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:scan_ -s 2 -c 1 -o $O/prof_scan_$TAG python tools/ncu_target.py --op scan --S 16 --dist cyclic --map intra --L 256 --N 2097152 --dtype i32 > $O/ncu_scan_$TAG.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:reduce_ -s 2 -c 1 -o $O/prof_reduce_$TAG python tools/ncu_target.py --op reduce --S 8 --dist block --map intra --L 64 > $O/ncu_reduce_$TAG.log 2>&1
if [ "$2" != "quick" ]; then
  timeout 600 python bench.py --oracle-timing $O/oracle_timing_$TAG.jsonl > $O/oracle_timing_$TAG.log 2>&1
  timeout 2400 python tools/sweep.py --out $O/sweep_$TAG.jsonl > $O/sweep_$TAG.log 2>&1; echo SWEEP_RC=$? >> $O/sweep_$TAG.log
  timeout 120 python tools/resource_table.py $TAG > /dev/null 2>&1
  # the driver's own command under the launch-list pass
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_full_$TAG.csv python bench.py > $O/bench_ncu_full_$TAG.log 2>&1
  for tool in memcheck racecheck synccheck; do
    extra=""; [ $tool != memcheck ] && extra="--no-dp"
    timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py $extra > $O/${tool}_$TAG.log 2>&1
    echo "RC=$?" >> $O/${tool}_$TAG.log
  done
fi
ls $O
