# A/B of the cyclic cluster scan exchange: cluster barrier (default) vs st.async pushes (CUDANP_SCL_PUSH=1)
O=gpurun_out; mkdir -p $O/sanitizer; P=paper_conf_ppopp_yangz14_b200
CUDANP_LIB=$P/libcudanp_push.so timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_property.py -m gpu -q -k cluster > $O/exp_push_test.log 2>&1; echo RC=$? >> $O/exp_push_test.log
CUDANP_LIB=$P/libcudanp_push.so timeout 600 compute-sanitizer --tool memcheck python tools/sanitize_cases.py --quick --no-dp > $O/sanitizer/memcheck_push.log 2>&1; echo RC=$? >> $O/sanitizer/memcheck_push.log
for rep in 1 2; do for v in base push; do
  LIB=$P/libcudanp.so; [ $v = push ] && LIB=$P/libcudanp_push.so
  CUDANP_BIG_OPS=scan timeout 300 python tools/sweep.py --configs BIG --lib $LIB --out $O/exp_push_${v}_$rep.jsonl > /dev/null 2>&1
done; done
CUDANP_LIB=$P/libcudanp_push.so timeout 600 compute-sanitizer --tool racecheck python tools/sanitize_cases.py --quick --no-dp > $O/sanitizer/racecheck_push.log 2>&1; echo RC=$? >> $O/sanitizer/racecheck_push.log
