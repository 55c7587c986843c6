for nz in 64 128 40; do
  for z in auto 32 16 8; do
    if [ $z = auto ]; then python tools/cg_slab_time.py 512 512 $nz; else NB_CG_ZC=$z python tools/cg_slab_time.py 512 512 $nz; fi
  done
done > gpurun_out/zc_model.log 2>/dev/null
for z in auto 32 16; do if [ $z = auto ]; then python tools/cg_slab_time.py 320 320 40; else NB_CG_ZC=$z python tools/cg_slab_time.py 320 320 40; fi; done >> gpurun_out/zc_model.log 2>/dev/null
for z in auto 32; do if [ $z = auto ]; then python tools/cg_slab_time.py 512 512 512 32; else NB_CG_ZC=$z python tools/cg_slab_time.py 512 512 512 32; fi; done >> gpurun_out/zc_model.log 2>/dev/null
