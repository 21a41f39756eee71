#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py -q -x -m gpu > gpurun_out/r4f_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r4f_pytest.log
tail -2 gpurun_out/r4f_pytest.log; grep -E "^FAILED|Error" gpurun_out/r4f_pytest.log | head -5
python - <<'P' > gpurun_out/r4f_ngram_parity.log 2>&1
# parity of the generated kernel with 64 / 128 trigram outputs (one group beyond 64) and Plan 2 vs the oracle
import sys, numpy as np, torch
sys.path.insert(0, '.')
from oracle import oracle
from paper_conf_asplos_wangwdz0d24_b200 import rap, synth
from tests.parity import assert_parity
for name, w in [("ngram64", synth.c2_terabyte(0, n_ngram=64)), ("ngram128", synth.c2_terabyte(0, n_ngram=128)), ("plan2", synth.plan_graph(2, 0))]:
    for B in (1000, 4099):
        h = synth.make_batch(w, B, seed=5)
        plan = rap.Plan(w.spec, device=0)
        raw = rap.DeviceBatch(h, "cuda:0"); out = rap.DeviceOutput(plan, B, raw.sp_nnz, "cuda:0")
        plan.preprocess(raw, out); torch.cuda.synchronize()
        info = plan.info()
        got = out.to_numpy(); want = oracle.run(w.spec, h)
        assert_parity(got, want)
        print(name, B, "kernel", info["kernel_last"], "groups", info["rb_feature_groups"], "OK")
        plan.close()
P
tail -8 gpurun_out/r4f_ngram_parity.log
timeout 900 python bench.py --steps 300 --warmup 10 --no-corun --no-fusion --no-cpu-baseline --no-e2e --no-c4 --ngram-sweep 8,64,128 > gpurun_out/r4f_bench.json 2> gpurun_out/r4f_bench.err; tail -3 gpurun_out/r4f_bench.err
python - <<'P'
import json
d=json.loads(open('gpurun_out/r4f_bench.json').read().strip().splitlines()[-1])
print('c2', d['ms_per_step'], d['roofline']['frac'])
for x in d['ngram_sweep']: print(x)
print('plans', [(p.get('workload'), p.get('kernel'), p.get('kernel_ms'), p.get('frac')) for p in d['plans']])
P
