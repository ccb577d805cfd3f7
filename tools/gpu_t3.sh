set -x
timeout 600 python -m pytest tests/test_trsm_panel_gpu.py -x -q 2>&1 | tail -5 > gpurun_out/t3_test.txt
for EX in 0 1; do
  BLAS3_PANEL_EXTRA=$EX timeout 300 python tools/opt_ab.py trsm_nb 2048 4096 8192 --cases strsm,strsm8k4k,strsm4096,strsm2048 --rounds 3 > gpurun_out/t3_ab_ex$EX.txt 2>&1
done
TL_OPTS='{"trsm_nb": 8192}' timeout 120 python tools/timeline.py strsm 8192 > gpurun_out/t3_tl8192.txt 2>&1
TL_OPTS='{"trsm_nb": 4096}' timeout 120 python tools/timeline.py strsm 8192 > gpurun_out/t3_tl4096.txt 2>&1
TL_OPTS='{"trsm_nb": 2048}' timeout 120 python tools/timeline.py strsm 8192 > gpurun_out/t3_tl2048.txt 2>&1
