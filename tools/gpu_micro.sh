set -x
cd tools/micro
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/simd16 simd16.cu && /tmp/simd16 > ../../gpurun_out/simd16.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lat lat.cu && /tmp/lat >> ../../gpurun_out/simd16.log 2>&1
cat ../../gpurun_out/simd16.log
