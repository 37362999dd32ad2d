# build a variant of the package with extra nvcc flags: tools/mkvariant.sh NAME "-DX=1 ..."
set -e
d=build_variants/$1
rm -rf $d && mkdir -p $d
cp -r paper_conf_dac_lugklr25_b200 include $d/
rm -rf $d/paper_conf_dac_lugklr25_b200/build $d/paper_conf_dac_lugklr25_b200/libinsta.so
(cd $d && INSTA_NVCC_EXTRA="$2" python -m paper_conf_dac_lugklr25_b200.build > /dev/null 2>&1)
ls -la $d/paper_conf_dac_lugklr25_b200/libinsta.so
