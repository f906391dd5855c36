# A/B of 3D kernel variants on one box: base lib vs new lib (clusters off / on); parity first
# usage: bash tools/ab3d.sh TAG
TAG=${1:-ab}
mkdir -p gpurun_out
export MRLBM_CLUSTER=2
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py -q -m gpu -k "D3Q or 3d" -x > gpurun_out/${TAG}_pytest_cl2.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_cl2.log
unset MRLBM_CLUSTER
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "D3Q" -x > gpurun_out/${TAG}_pytest_cl1.log 2>&1; tail -2 gpurun_out/${TAG}_pytest_cl1.log
for rep in 1 2; do
for cfg in "C3 fp64" "C5 fp64" "C4 fp32"; do set -- $cfg
  MRLBM_LIB=$PWD/ab/libmrlbm_base.so timeout 300 python bench.py --config $1 --precision $2 --steps 200 --no-cpu-baseline | sed 's/^{/{"lib": "base", /' >> gpurun_out/${TAG}.jsonl
  MRLBM_CLUSTER=1 timeout 300 python bench.py --config $1 --precision $2 --steps 200 --no-cpu-baseline | sed 's/^{/{"lib": "new_cl1", /' >> gpurun_out/${TAG}.jsonl
  MRLBM_CLUSTER=2 timeout 300 python bench.py --config $1 --precision $2 --steps 200 --no-cpu-baseline | sed 's/^{/{"lib": "new_cl2", /' >> gpurun_out/${TAG}.jsonl
done
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
