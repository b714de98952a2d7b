#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small GPU parity cases.
set -u
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py tests/test_nbody.py tests/test_gpu_edge.py tests/test_gpu_r2.py -m gpu -q -x \
      -k "test_stream_bit_exact and 3-2-4 or test_hotspot_bit_exact and 3-4-shape0 or test_hotspot_temporal_block_bit_exact and 3-1-shape1-8 or test_stencil_reduction and 3 or test_sgemm and 1-2-shape0 or test_cholesky_exact_factor and 2-5-nb1 or test_cholesky_exact_factor and 1-4-nb2 or test_blackscholes and 2-4 or test_nbody_gpu_vs_oracle or test_sgemm_dp_chunks and 4-shape0 or test_sgemm_splitk or test_stream_tiny and 3-3-5 or test_hotspot_degenerate_grids and 3-4-shape1 or test_sgemm and 2-1-shape2 or test_sgemm and 2-1-shape3 or test_graph_recaptured or test_green_context_dp_perf or test_green_context_caller_stream" \
      > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"
  grep -E "ERROR SUMMARY|passed|failed" gpurun_out/sanitize_$tool.log | tail -3
done
