timeout 900 python -m pytest tests/test_trsm_panel_gpu.py tests/test_trsm_sweep_gpu.py tests/test_graph_gpu.py -x -q 2>&1 | tail -3 > gpurun_out/t6_test.txt
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_parity_large_gpu.py -x -q -k "strsm or trsm" 2>&1 | tail -3 >> gpurun_out/t6_test.txt
for f in 0 20; do for p in 0 1; do
  echo "FREE=$f PANEL2=$p" >> gpurun_out/t6_tl.txt
  BLAS3_PANEL2_FREE=$f TL_OPTS="{\"trsm_panel2\": $p}" timeout 120 python tools/timeline.py strsm 8192 2>&1 | grep -v arn >> gpurun_out/t6_tl.txt
done; done
timeout 600 python tools/sustained_ab.py --rounds 3 sgemm strsm:trsm_panel2=0 strsm:trsm_panel2=1 > gpurun_out/t6_ab.txt 2>&1
BLAS3_PANEL2_FREE=20 timeout 600 python tools/sustained_ab.py --rounds 3 sgemm strsm:trsm_panel2=0 strsm:trsm_panel2=1 > gpurun_out/t6_ab20.txt 2>&1
timeout 300 python tools/opt_ab.py trsm_panel2 0 1 --cases strsm,strsm4096,strsm2048,strsm8k4k --rounds 3 > gpurun_out/t6_opt.txt 2>&1
