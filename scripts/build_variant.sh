# usage: build_variant.sh OUT.so -DFLAG=.. ...   (both translation units of libdyc.so, one nvcc call)
out=$1; shift
nvcc -O3 -std=c++17 -lineinfo -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -shared -cudart static -ldl \
  -I include "$@" -o $out paper_conf_icde_lizlhs21_b200/csrc/dyc_api.cu paper_conf_icde_lizlhs21_b200/csrc/dyc_dist.cu
