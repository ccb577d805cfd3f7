"""Static SASS size of each kernel attributed to source lines (uses the
-lineinfo tables): python tools/sass_size.py [kernel-substring] [top]"""
import collections, os, re, subprocess, sys, tempfile

so = os.path.join(os.path.dirname(__file__), "..", "paper_conf_ipps_cuiwxyf11_b200", "libblas3.so")
want = sys.argv[1] if len(sys.argv) > 1 else "tc_structured_gemmILi1"
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
with tempfile.TemporaryDirectory() as d:
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(so)], cwd=d, capture_output=True)
    out = ""
    for f in os.listdir(d):
        out += subprocess.run(["nvdisasm", "-gi", os.path.join(d, f)], capture_output=True, text=True).stdout
fn, loc = None, None
cnt = collections.Counter()
for line in out.splitlines():
    m = re.match(r"\s*\.text\.(\S+):", line) or re.match(r"(\S+):\s*$", line)
    if m and "_Z" in m.group(1):
        fn = m.group(1)
    m = re.search(r'//## File "([^"]+)", line (\d+)', line)
    if m:
        loc = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    if fn and want in fn and re.search(r"/\*[0-9a-f]{4,6}\*/\s+[A-Z@]", line):
        cnt[loc] += 1
tot = sum(cnt.values())
print(f"{want}: {tot} instructions ({tot * 16 / 1024:.1f} KB)")
for (f, l), c in cnt.most_common(top):
    print(f"  {f}:{l:<5d} {c:6d}")
