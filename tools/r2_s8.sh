# round-2 session 8: 2D 6-deep ring defaults: tests, bench, ncu; C4 ring A/B
mkdir -p gpurun_out
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s8_smoke.log 2>&1 || { echo smoke failed; exit 1; }
timeout 1200 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/r2s8_pytest.log 2>&1; tail -2 gpurun_out/r2s8_pytest.log
timeout 600 python bench.py > gpurun_out/r2s8_default.json 2> gpurun_out/r2s8_default.err
timeout 300 python bench.py --steps 20 --warmup 3 > gpurun_out/r2s8_k20.json 2> gpurun_out/r2s8_k20.err
timeout 300 python bench.py --config C2 --precision fp32 > gpurun_out/r2s8_c2fp32.json 2> gpurun_out/r2s8_c2fp32.err
python tools/show_bench.py gpurun_out/r2s8_default.json gpurun_out/r2s8_k20.json gpurun_out/r2s8_c2fp32.json
for rep in 1 2; do
  timeout 200 python bench.py --config C4 --steps 200 --no-cpu-baseline --no-e2e | sed 's/^{/{"lib": "S4", /' >> gpurun_out/r2s8_c4ring.jsonl
  MRLBM_TILE=3 timeout 200 python bench.py --config C4 --steps 200 --no-cpu-baseline --no-e2e | sed 's/^{/{"lib": "S6", /' >> gpurun_out/r2s8_c4ring.jsonl
done
python tools/show_ab.py gpurun_out/r2s8_c4ring.jsonl
bash tools/ncu_capture.sh r02s8 "C2 fp64" "C2 fp32" > /dev/null 2>&1
ls gpurun_out | grep r02s8 | head
