mkdir -p gpurun_out/stv
for v in zc4m8 zc2m16 zc4m12 zc2m12 rint; do
  TACKER_LIB=$PWD/varlibs/lib_$v.so timeout 300 python tools/be_table.py stencil,mriq,mrifhd > gpurun_out/stv/$v.json 2>&1
done
