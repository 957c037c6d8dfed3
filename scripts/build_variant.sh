# build an experimental library variant: build_variant.sh <name> <nvcc defines...>
#   -> paper_conf_ipps_juryl022_b200/lib/exp_<name>/libmstamp_b200.so (CSRC=<dir> to build another source tree)
set -e
name=$1; shift
out=$PWD/paper_conf_ipps_juryl022_b200/lib/exp_$name
mkdir -p $out/obj
C=${CSRC:-paper_conf_ipps_juryl022_b200/csrc}
INC=${INC:-$PWD/include}
export out INC
(cd $C && ls mp_kernels.cu mp_seed_tc.cu mp_api.cpp inst_*.cu) | xargs -P $(nproc) -I{} sh -c \
  "nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC -I $INC $* -c $C/{} -o $out/obj/{}.o || echo FAILED {}"
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $out/libmstamp_b200.so $out/obj/*.o -lcudart
rm -rf $out/obj
