# A/B round 2c: per-row mbarrier exchange (new default) vs CTA-wide barrier (ab/libmrlbm_ctabar.so)
TAG=${1:-ab}
mkdir -p gpurun_out
timeout 90 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { echo "smoke failed/hung"; tail -5 gpurun_out/${TAG}_smoke.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_p2p.py tests/test_gpu_slabs.py -q -m gpu -x -k "D3Q or 3d or p2p or slab" --timeout 120 > gpurun_out/${TAG}_pytest.log 2>&1; tail -2 gpurun_out/${TAG}_pytest.log
timeout 600 python -m pytest tests/test_gpu_parity_long.py -q -m gpu -x -k "3d" --timeout 200 > gpurun_out/${TAG}_pytest_long.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_long.log
run() { local tag=$1; shift
  env "$@" timeout 150 python bench.py --steps 200 --no-cpu-baseline $BARGS | sed "s/^{/{\"lib\": \"$tag\", /" >> gpurun_out/${TAG}.jsonl; }
for rep in 1 2; do
  for B in "--config C3" "--config C5" "--config C4"; do BARGS="$B"
    run rowbar X=1; run ctabar MRLBM_LIB=$PWD/ab/libmrlbm_ctabar.so
  done
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
