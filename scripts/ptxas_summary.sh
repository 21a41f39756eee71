#!/bin/bash
# ptxas register / spill summary of librap's kernels (dev tool)
python -m paper_conf_asplos_wangwdz0d24_b200._build 2>&1 | python3 -c "
import sys,re
fn=None
for ln in sys.stdin:
    m=re.search(r'Function properties for (\S+)', ln)
    if m: fn=m.group(1); continue
    m=re.search(r'(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads', ln)
    if m and fn and '${1:-Li32ELi64}' in fn:
        n=re.sub(r'^_ZN4rapk\d+','',fn)[:48]
        print(f'{n:50s} frame {m.group(1):>5s} st {m.group(2):>5s} ld {m.group(3):>5s}')
    m=re.search(r'Used (\d+) registers', ln)
"
