# build an experimental library variant into /tmp-like dir under the repo: build_variant.sh <name> <nvcc defines...>
set -e
name=$1; shift
out=paper_conf_ipps_juryl022_b200/lib/exp_$name
mkdir -p $out/obj
C=paper_conf_ipps_juryl022_b200/csrc
for f in mp_kernels.cu mp_api.cpp $(cd $C && ls inst_*.cu); do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC -I include "$@" -c $C/$f -o $out/obj/$f.o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $out/libmstamp_b200.so $out/obj/*.o -lcudart
rm -rf $out/obj
