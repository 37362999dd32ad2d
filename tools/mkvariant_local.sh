# Build a variant of libinsta.so HERE (cross-compile) with extra nvcc flags for one source file,
# relinking with the default build's objects: tools/mkvariant_local.sh NAME SOURCE "-DX=1 ..."
set -e
d=build_variants/$1; src=$2; flags=$3
rm -rf $d && mkdir -p $d/obj
cp -r paper_conf_dac_lugklr25_b200 include tools $d/
rm -rf $d/paper_conf_dac_lugklr25_b200/build
objs=""
for o in paper_conf_dac_lugklr25_b200/build/*.o; do
  b=$(basename $o .o)
  if [ "$b" = "$src" ]; then
    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --fmad=false -lineinfo -Xcompiler -fPIC $flags -I include -c paper_conf_dac_lugklr25_b200/csrc/$src -o $d/obj/$b.o
    objs="$objs $d/obj/$b.o"
  else
    objs="$objs $o"
  fi
done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $d/paper_conf_dac_lugklr25_b200/libinsta.so $objs -cudart static
touch -c $d/paper_conf_dac_lugklr25_b200/libinsta.so
