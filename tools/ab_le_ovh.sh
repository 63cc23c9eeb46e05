# A/B of the LE inter-warp register budget (CUDANP_LE_INTER_OVH 56 default vs 40)
O=gpurun_out; mkdir -p $O; P=paper_conf_ppopp_yangz14_b200
timeout 600 python -m pytest tests/test_gpu_le.py -m gpu -q > $O/exp_leovh_test_56.log 2>&1; echo RC=$? >> $O/exp_leovh_test_56.log
for rep in 1 2; do
  timeout 900 python tools/sweep.py --configs F2 --lib $P/libcudanp.so --out $O/exp_leovh_56_$rep.jsonl > /dev/null 2>&1
  timeout 900 python tools/sweep.py --configs F2 --lib $P/libcudanp_ovh40.so --out $O/exp_leovh_40_$rep.jsonl > /dev/null 2>&1
done
