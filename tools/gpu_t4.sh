for cfg in "0 0" "1 0" "1 1" "1 2" "1 4"; do set -- $cfg
  echo "EX=$1 XW=$2" >> gpurun_out/t4.txt
  for nb in 8192 2048; do
    BLAS3_TRSM_NB=$nb BLAS3_PANEL_EXTRA=$1 BLAS3_PANEL_XW=$2 timeout 120 python tools/timeline.py strsm 8192 2>&1 | grep -E 'panel_kernel|span' >> gpurun_out/t4.txt
  done
done
BLAS3_TRSM_NB=8192 BLAS3_PANEL_EXTRA=1 BLAS3_TRACE_PANEL=1 timeout 120 python tools/strsm_once.py 8192 > gpurun_out/t4_trace_ex1.txt 2>&1
BLAS3_TRSM_NB=8192 BLAS3_PANEL_EXTRA=0 BLAS3_TRACE_PANEL=1 timeout 120 python tools/strsm_once.py 8192 > gpurun_out/t4_trace_ex0.txt 2>&1
