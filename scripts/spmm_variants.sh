#!/bin/bash
# SpMM library variants: integer-exact parity subset + per-config spmm loop time (interleaved, 2 rounds).
# usage: gpurun -- 'bash scripts/spmm_variants.sh TAG lib1.so lib2.so ...' (libs under the package dir)
TAG=$1; shift
mkdir -p gpurun_out
for lib in "$@"; do
  LF_LIB=$PWD/paper_conf_hpdc_pengtpk25_b200/$lib timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x \
     -k "integer_exact or full_config or full_reddit" > gpurun_out/${TAG}_${lib}_pytest.txt 2>&1
  echo "$lib $(tail -1 gpurun_out/${TAG}_${lib}_pytest.txt)" >> gpurun_out/${TAG}_summary.txt
done
for rep in 1 2; do
for c in ${CFGS:-c2_rmat20 c3_stencil126 c4_reddit}; do
  for lib in "$@"; do
    r=$(LF_LIB=$PWD/paper_conf_hpdc_pengtpk25_b200/$lib timeout 300 python scripts/spmm_time.py $c iters=20 | tail -1)
    echo "$rep $lib $c $(echo "$r" | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["spmm_loop_ms"], d["params"]["n_parts"])')" >> gpurun_out/${TAG}_summary.txt
  done
done
done
cat gpurun_out/${TAG}_summary.txt
