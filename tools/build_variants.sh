# Build library variants for an A/B run: tools/build_variants.sh name:"-DFLAG=1 ..." ...
# -> paper_conf_sigmod_paullhl21_b200/libmgj_<name>.so (run them with tools/gpu_ab2.sh)
R=$(cd "$(dirname "$0")/.." && pwd)
for v in "$@"; do
  n=${v%%:*}; f=${v#*:}
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -shared -I "$R/include" $f \
    -o "$R/paper_conf_sigmod_paullhl21_b200/libmgj_$n.so" "$R/paper_conf_sigmod_paullhl21_b200/csrc/mgj.cu" &
done
wait
