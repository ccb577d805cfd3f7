"""Summarise ncu outputs into profiles/ (committed evidence).

usage: python tools/ncu_summary.py <tag> <launches.csv> <prof.ncu-rep> [flops_per_launch]
writes profiles/<tag>_launches.md, profiles/<tag>_sgemm_ncu.md, profiles/ncu_sgemm_traffic.json
"""
import collections, csv, json, os, subprocess, sys

tag, launches, rep = sys.argv[1], sys.argv[2], sys.argv[3]
flops = float(sys.argv[4]) if len(sys.argv) > 4 else 2.0 * 8192 ** 3
os.makedirs("profiles", exist_ok=True)

# ---- launch list (one bench step, serialized & cold under ncu: compare shares)
rows = list(csv.reader(open(launches)))
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hi]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
seq = [(r[ki].split("(")[0], float(r[vi].replace(",", "")) / 1e6) for r in rows[hi + 1:] if len(r) > vi]
tot = sum(t for _, t in seq)
agg = collections.OrderedDict()
for n, t in seq:
    a = agg.setdefault(n, [0, 0.0]); a[0] += 1; a[1] += t
routine_bounds = []  # first 5 tc launches = sgemm, ssymm, ssyrk, ssyr2k, strmm
with open(f"profiles/{tag}_launches.md", "w") as f:
    f.write(f"# {tag}: kernel launch list of one bench step (ncu gpu__time_duration, "
            f"--clock-control none; serialized, cold caches: compare shares, not absolutes)\n\n")
    f.write(f"command: `ncu --metrics gpu__time_duration.sum --clock-control none python bench.py "
            f"--steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-alt-mode --no-context --no-routine-clocks`\n\n")
    f.write(f"total kernel time {tot:.3f} ms over {len(seq)} launches\n\n")
    f.write("| kernel | launches | total ms | share |\n|---|---|---|---|\n")
    for n, (c, t) in agg.items():
        f.write(f"| {n} | {c} | {t:.3f} | {100*t/tot:.1f}% |\n")
    f.write("\nfirst launches in order (ms): the chain sgemm, ssymm, ssyrk, ssyr2k, strmm(+copy), strsm(...)\n\n")
    for n, t in seq[:12]:
        f.write(f"- {n}: {t:.3f}\n")

# ---- full capture of the sgemm launch
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
H, U, V = r[0], r[1], r[2]
def get(name):
    for i, n in enumerate(H):
        if n == name:
            return V[i], U[i]
    return None, None
keys = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__ops_path_tensor_op_utchmma_src_tf32_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum",
        "l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__mem_tensor_reads_op_utcmma_matrix_c.sum.pct_of_peak_sustained_elapsed",
        "smsp__mem_tensor_writes_op_utcmma.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__sass_inst_executed_op_utcmma.sum",
        "smsp__sass_inst_executed_op_global_st.sum", "smsp__sass_inst_executed_op_global_ld.sum",
        "smsp__sass_inst_executed_op_shared_st.sum", "smsp__sass_inst_executed_op_shared_ld.sum",
        "smsp__inst_executed_op_ldgsts.sum", "lts__t_sectors_srcunit_tex_op_write.sum"]
vals = {}
for k in keys:
    v, u = get(k)
    if v is not None:
        vals[k] = (v, u)
def num(k, scale=1.0):
    v, u = vals.get(k, (None, None))
    if v is None:
        return None
    x = float(v.replace(",", ""))
    mult = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "nsecond": 1e-9, "usecond": 1e-6,
            "msecond": 1e-3, "second": 1.0, "ms": 1e-3, "us": 1e-6, "ns": 1e-9}.get(u, 1.0)
    return x * mult * scale
dur = num("gpu__time_duration.sum")
rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
traffic = (rd or 0) + (wr or 0)
alg_bytes = 3 * 8192 * 8192 * 4 + 8192 * 8192 * 4   # A, B, C read once, C written once
with open(f"profiles/{tag}_sgemm_ncu.md", "w") as f:
    f.write(f"# {tag}: ncu --set full of tc_structured_gemm (SGEMM NN, N=8192, alpha=1.5, beta=0.5)\n\n")
    f.write("command: `ncu --set full --clock-control none --import-source on -k regex:tc_structured "
            "-c 1 python tools/one_call.py sgemm 8192`\n\n")
    f.write("| metric | value | unit |\n|---|---|---|\n")
    for k, (v, u) in vals.items():
        f.write(f"| {k} | {v} | {u} |\n")
    if dur:
        f.write(f"\nunder ncu: {flops/dur/1e12:.1f} TF/s algorithmic (2N^3 / duration)\n")
    f.write(f"\nDRAM traffic per launch: {traffic/1e6:.1f} MB vs algorithmic minimum "
            f"{alg_bytes/1e6:.1f} MB (A, B, C read once + C written once) -> "
            f"{traffic/alg_bytes:.2f}x\n")
stamp = os.path.join("paper_conf_ipps_cuiwxyf11_b200", "libblas3.so.sha256")
lib_sha = open(stamp).read().strip() if os.path.exists(stamp) else None
json.dump({"tag": tag, "kernel": "tc_structured_gemm (sgemm NN N=8192)",
           "dram_bytes_per_launch": traffic, "dram_read": rd, "dram_write": wr,
           "algorithmic_bytes": alg_bytes, "source": f"profiles/{tag}_sgemm_ncu.md",
           "lib_sha256": lib_sha},
          open("profiles/ncu_sgemm_traffic.json", "w"), indent=1)
print(open(f"profiles/{tag}_launches.md").read())
print(open(f"profiles/{tag}_sgemm_ncu.md").read())
