#!/bin/bash
# quick iteration: build, gpu tests, probe, trace (dev tool)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests -x -q -m gpu 2>&1 | tail -4
timeout 300 python scripts/probe.py
timeout 120 python scripts/trace.py
