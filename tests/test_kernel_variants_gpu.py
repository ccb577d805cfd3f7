"""The opt-in kernel variants selected by environment variables at library
load (they are cached once per process, hence subprocesses): the CTA-pair
tcgen05 kernel (BLAS3_TC_CTA=2, cta_group::2) and the static tile schedule
(BLAS3_TC_STATIC=1), the single-CTA kernel (BLAS3_TC_CTA=1; the default
picks the pair kernel for large problems), whole tiles only
(BLAS3_TC_SPLIT=0: no k-sliced tail), and the GM_map adaptor forced on at
every size (BLAS3_GM_MAP=1: transposed / symmetric / triangular operands
materialised in global memory first, the default only for large problems), and
STRSM's first panel by update + solve instead of the precomputed Y - M X form
(BLAS3_TRSM_FIRST_YM=0), the per-thread 4-B epilogue accesses of C instead of
the 16-B vector ones (BLAS3_TC_VEC_STORE=0) and no L2 prefetch of C
(BLAS3_TC_C_PREFETCH=0), C read by cp.async two groups ahead into shared memory
instead of one group ahead in registers (BLAS3_TC_C_ASYNC=1), and 16 k-blocks per TMEM partial
(BLAS3_TC_KC=16: only the bit-exact integer pins run there -- its rounding
error exceeds the fp32-class diagnostic by design, Q24).  Each child
process runs a representative subset of the parity suite (every routine
family, both transposes/sides) on that variant."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("env", [{"BLAS3_TC_CTA": "1"}, {"BLAS3_TC_CTA": "2"}, {"BLAS3_TC_STATIC": "1"},
                                 {"BLAS3_TC_SPLIT": "0"}, {"BLAS3_TC_CTA": "1", "BLAS3_TC_SPLIT": "0"},
                                 {"BLAS3_GM_MAP": "1"}, {"BLAS3_TRSM_FIRST_YM": "0"},
                                 {"BLAS3_TC_VEC_STORE": "0", "BLAS3_TC_C_PREFETCH": "0"}, {"BLAS3_TC_KC": "16"},
                                 {"BLAS3_TC_C_ASYNC": "1"}],
                         ids=["single_cta", "cta_pair", "static_schedule", "no_split", "single_cta_no_split",
                              "gm_map", "trsm_no_first_ym", "scalar_epilogue", "kc16", "c_by_cp_async"])
def test_variant_subset(env):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    sel = "3xtf32 and (sgemm or ssymm or syrk or strmm or strsm or split_is_real)"
    if env.get("BLAS3_TC_KC") == "16":
        sel = "3xtf32 and (integer or split_is_real)"      # bit-exact pins: independent of the chunk
    cmd = [sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-k", sel,
           os.path.join(ROOT, "tests", "test_parity_gpu.py")]
    r = subprocess.run(cmd, env={**os.environ, **env}, cwd=ROOT, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout
