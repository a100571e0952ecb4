#!/bin/bash
# compute-sanitizer passes over small GPU parity cases.
mkdir -p gpurun_out
SEL="test_query_batch_bit_exact or test_reuse_and_modes_bit_exact or test_edge_queries or test_decode_list_roundtrip or test_intersect_sets_match_oracle or test_docid_sharding or test_decode_edge_lists or test_entry_budget or test_large_tf or test_peer_exchange_shards_on_one_device or test_decode_all_checksum"
for tool in memcheck racecheck synccheck; do
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi.py -q -x -k "$SEL" > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_$tool.log | tail -2 | tr '\n' ' ')"
done
