cd /root/repo
MM_TRSM_COL=0 timeout 1200 compute-sanitizer --tool racecheck --error-exitcode 9 --print-limit 5 \
    python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "test_cholesky_exact_factor and 2-5-nb1" > gpurun_out/san_rc0.log 2>&1
echo "col0 rc=$?"; grep -c "Race reported" gpurun_out/san_rc0.log; grep -m2 "Race reported" gpurun_out/san_rc0.log | cut -c1-150
MM_GEMM_PAIR=0 timeout 1200 compute-sanitizer --tool racecheck --error-exitcode 9 --print-limit 5 \
    python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "test_cholesky_exact_factor and 2-5-nb1 or test_cholesky_random_spd and nb1" > gpurun_out/san_rc1.log 2>&1
echo "nopair rc=$?"; grep -c "Race reported" gpurun_out/san_rc1.log; grep -E "passed|failed" gpurun_out/san_rc1.log
