# which build keeps the slab / P2P results bitwise equal to one rank: in-tree (rotated), -fmad=false, no rotation
for lib in cur nofmad norot; do
  if [ "$lib" = cur ]; then L=""; else L=$PWD/ab/libmrlbm_$lib.so; fi
  MRLBM_LIB=$L timeout 600 python -m pytest tests/test_gpu_slabs.py tests/test_gpu_p2p.py -m gpu -q > gpurun_out/bitwise_$lib.log 2>&1; echo "$lib: $(tail -n 1 gpurun_out/bitwise_$lib.log)"
done
bash tools/ab_libs.sh ab12 "cur nofmad norot" "C5 fp64" "C3 fp64"
