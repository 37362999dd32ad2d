# cone-pass probe (default build and INSTA_SL_PHASES variant) + Top-K sigma parity with the propagated taint
mkdir -p gpurun_out/cone /tmp/tr
timeout 900 python -m pytest tests/test_gpu_topk.py -q -k "sigma_parity" > gpurun_out/cone/topk.log 2>&1; echo "topk rc=$?" >> gpurun_out/cone/topk.log
tail -3 gpurun_out/cone/topk.log
timeout 600 python tools/cone_probe.py C4 1e-7 1e-6 1e-5 1e-4 > gpurun_out/cone/c4.log 2>&1; echo "c4 rc=$?"
timeout 600 python tools/cone_probe.py C3 1e-6 1e-4 1e-3 1e-2 > gpurun_out/cone/c3.log 2>&1; echo "c3 rc=$?"
cd build_variants/phases
INSTA_SL_TRACE=/tmp/tr timeout 600 python tools/cone_probe.py C3 1e-4 1e-2 > ../../gpurun_out/cone/c3_phases.log 2>&1; echo "c3p rc=$?"
INSTA_SL_TRACE=/tmp/tr timeout 600 python tools/cone_probe.py C4 1e-7 1e-5 > ../../gpurun_out/cone/c4_phases.log 2>&1; echo "c4p rc=$?"
