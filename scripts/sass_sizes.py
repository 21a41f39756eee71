#!/usr/bin/env python
"""SASS instruction count per source function of the fused kernel (dev tool)."""
import collections, os, re, subprocess, sys, tempfile
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
lib = os.path.join(ROOT, "paper_conf_asplos_wangwdz0d24_b200", "librap.so")
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=d, capture_output=True)
cub = max((os.path.join(d, f) for f in os.listdir(d) if f.endswith(".cubin")), key=os.path.getsize)
txt = subprocess.run(["nvdisasm", "--print-line-info", cub], capture_output=True, text=True).stdout
src = open(os.path.join(ROOT, "paper_conf_asplos_wangwdz0d24_b200", "csrc", "rap_kernel.cu")).read().split("\n")
starts = [(i, m.group(1)) for i, l in enumerate(src, 1) if (m := re.match(r"(?:__device__|__global__)[^(]*?(\w+)\(", l))]
cur = sec = None
cnt = collections.Counter()
for ln in txt.splitlines():
    if ln.lstrip().startswith(".section") and ".text." in ln:
        sec = ln
    m = re.search(r'"([^"]+)", line (\d+)', ln)
    if m:
        f = m.group(1).split("/")[-1]
        cur = int(m.group(2)) if f == "rap_kernel.cu" else f
        continue
    if re.match(r"\s+/\*[0-9a-f]{4,}\*/", ln) and sec and "32ELi64" in sec:
        cnt[cur] += 1
agg = collections.Counter()
for k, v in cnt.items():
    name = k if not isinstance(k, int) else max(((i, n) for i, n in starts if i <= k), default=(0, "?"))[1]
    agg[name] += v
for k, v in agg.most_common(int(sys.argv[1]) if len(sys.argv) > 1 else 20):
    print(v, k)
print("total", sum(cnt.values()))
