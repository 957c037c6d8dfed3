# build an experimental library variant: build_variant.sh <name> <nvcc defines...>
#   -> paper_conf_ipps_juryl022_b200/lib/exp_<name>/libmstamp_b200.so
set -e
name=$1; shift
out=$PWD/paper_conf_ipps_juryl022_b200/lib/exp_$name
mkdir -p $out/obj $out/gen
C=$PWD/paper_conf_ipps_juryl022_b200/csrc
INC=$PWD/include
python -c "import sys; sys.path.insert(0, '$PWD'); from paper_conf_ipps_juryl022_b200 import build; build.generate_units('$out/gen')"
export out INC C
( (cd $C && ls mp_kernels.cu mp_seed_tc.cu mp_api.cpp | sed "s|^|$C/|"); ls $out/gen/*.cu ) | xargs -P $(nproc) -I{} sh -c \
  "nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC -I $INC -I $C $* -c {} -o $out/obj/\$(basename {}).o || echo FAILED {}"
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $out/libmstamp_b200.so $out/obj/*.o -lcudart
rm -rf $out/obj $out/gen
