for r in 1 2 3; do for d in 0 8192; do
  echo "DBG=$d round $r" >> gpurun_out/t16.txt
  BLAS3_DEBUG_TC=$d timeout 200 python tools/opt_ab.py pdl 1 --rounds 2 --cases sgemm,strsm,strmm,ts_syrk,ts_syr2k,sgemm2048,strsm4096 >> gpurun_out/t16.txt 2>&1
done; done
timeout 300 python tools/leaf_probe.py --rounds 3 > gpurun_out/t16_leaf.txt 2>&1
timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_split_tail_gpu.py tests/test_graph_gpu.py -q -x 2>&1 | tail -2 > gpurun_out/t16_test.txt
