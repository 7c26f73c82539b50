#!/bin/bash
# stream binding fix: e2e probe, bench C2 / C3, full GPU suite
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/e2e_probe.py C2 6 > gpurun_out/s3o_e2e_C2.txt 2>&1
timeout 900 python tools/e2e_probe.py C3 3 > gpurun_out/s3o_e2e_C3.txt 2>&1
timeout 900 python bench.py --no-cpu > gpurun_out/s3o_bench_C2.log 2>&1
timeout 1200 python bench.py --config C3 --no-cpu --no-gmres > gpurun_out/s3o_bench_C3.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/s3o_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/s3o_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3o_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/s3o_smoke.log
