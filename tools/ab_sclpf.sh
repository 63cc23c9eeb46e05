O=gpurun_out; mkdir -p $O
P=paper_conf_ppopp_yangz14_b200
for v in base pf1 pf2; do
  case $v in base) LIB=$P/libcudanp.so;; pf1) LIB=$P/libcudanp_sclpf1.so;; pf2) LIB=$P/libcudanp_sclpf2.so;; esac
  CUDANP_LIB=$LIB timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_property.py -m gpu -q -k "cluster" > $O/exp_sclpf_test_$v.log 2>&1; echo RC=$? >> $O/exp_sclpf_test_$v.log
done
for rep in 1 2; do for v in base pf1 pf2; do
  case $v in base) LIB=$P/libcudanp.so;; pf1) LIB=$P/libcudanp_sclpf1.so;; pf2) LIB=$P/libcudanp_sclpf2.so;; esac
  CUDANP_BIG_OPS=scan timeout 600 python tools/sweep.py --configs BIG --lib $LIB --out $O/exp_sclpf_${v}_$rep.jsonl > $O/exp_sclpf_sweep_${v}_$rep.log 2>&1
done; done
