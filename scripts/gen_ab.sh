#!/bin/bash
# A/B of generator builds: GEN_LIBS="abtest/lib_a.so ..." GEN_CFGS="c2 c4" [GEN_ENV="X=1"]
for rep in 1 2; do for lib in $GEN_LIBS; do
  echo "== $lib"; env MAGIS_LIB=$lib $GEN_ENV timeout 600 python scripts/gen_time.py ${GEN_CFGS:-c2 c5 c3 c4} 2>&1 | grep device
done; done
