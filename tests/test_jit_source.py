"""The code generator (rap_jit.cpp) without a GPU: for the config graphs and
random graphs, rap_debug_jit_source emits CUDA source that NVRTC compiles for
sm_100a, every sparse output gets its own straight-line block, and the
parameters appear as immediates.  Parity of the generated
kernel against the oracle is in tests/test_gpu_parity.py (kernel "jit")."""
import numpy as np
import pytest

from paper_conf_asplos_wangwdz0d24_b200 import synth
from tests.helpers import node, spec


@pytest.fixture(scope="module")
def rap():
    from paper_conf_asplos_wangwdz0d24_b200 import _build, rap as r

    _build.build()
    r.load()
    return r


def test_c2_source_compiles_with_immediates(rap):
    w = synth.c2_terabyte(0)
    st, src, ok, log = rap.jit_source(w.spec, compile=True)
    assert st == "OK" and ok, log
    # the batched emitter (rap_jit.cpp emit_batched): every output of the
    # plan in exactly one batch, in batches of at most 8
    import re

    listed = [int(f) for b in re.findall(r"// batch of outputs([ 0-9]+)", src) for f in b.split()]
    # every output in a batch; the dense-warp tail's outputs twice (the sparse
    # warps' copy for multi-chunk blocks, and emit_tail)
    assert sorted(set(listed)) == list(range(34)) and max(listed.count(f) for f in set(listed)) <= 2
    assert "kTail = true" in src
    assert all(len(b.split()) <= 8 for b in re.findall(r"// batch of outputs([ 0-9]+)", src))
    # the trigram outputs read their memoised sources from registers: 3 per
    # trigram emission (8 trigrams, plus any the dense-warp tail re-emits)
    n_m = src.count("(uint64_t)m")
    assert n_m >= 24 and n_m % 3 == 0
    # every SigridHash salt is an immediate H(salt) (R3)
    from oracle import oracle

    for nd in w.spec["nodes"]:
        if nd["op"] == "sigridhash":
            assert f"{oracle.H(nd['salt'])}ULL" in src


def test_c1_source_compiles(rap):
    w = synth.c1_kaggle(0)
    st, src, ok, log = rap.jit_source(w.spec, compile=True)
    assert st == "OK" and ok, log
    import re

    listed = [int(f) for b in re.findall(r"// batch of outputs([ 0-9]+)", src) for f in b.split()]
    assert sorted(set(listed)) == list(range(26)) and max(listed.count(f) for f in set(listed)) <= 2


@pytest.mark.parametrize("seed", range(3))
def test_random_graph_sources_compile(rap, seed):
    from tests.test_gpu_parity import _random_graph

    s = _random_graph(np.random.default_rng(100 + seed), 3, 4)
    st, src, ok, log = rap.jit_source(s, compile=True)
    assert st == "OK" and ok, log


def test_unsupported_plan(rap):
    nodes = [node("sigridhash", [("s", c)], salt=c, max_value=100) for c in range(70)]
    st, src, ok, log = rap.jit_source(spec(0, 70, nodes, list(range(70))), compile=False)
    assert st == "UNSUPPORTED"


def test_dense_chain_beyond_staged_ops(rap):
    """A dense chain of 101 ops exceeds what a DProg stages (kMaxDenseOps):
    its unit refers to the plan's global op pool (DUnit::gops), and the
    generated code must take those ops, not the DProg's staged array."""
    nodes, cur = [], ("d", 0)
    for i in range(100):
        nodes.append(node("fillnull", [cur], f_fill=0.125 * (i % 5)))
        cur = ("n", len(nodes) - 1)
    nodes.append(node("logit", [cur], eps=1e-3))
    nodes.append(node("sigridhash", [("s", 0)], salt=1, max_value=100))
    st, src, ok, log = rap.jit_source(spec(1, 1, nodes, [100, 101]), compile=False)
    assert st == "OK", log
    assert src.count("if (isnan(v)) v = ") == 100
    assert src.count("v = logf(__fdiv_rn(z, __fsub_rn(1.0f, z)))") == 1
    assert "expm1f" not in src  # no BoxCox in the graph
