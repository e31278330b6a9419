#!/bin/bash
# tools/mkvariant_rev.sh NAME REV  -> _vNAME/: the working tree with csrc/ at git revision REV, built
# (A/B of the working tree against a committed version: tools/ab.sh .,_vNAME WORKLOAD...)
set -e
N=$1; R=$2
D=_v$N
rm -rf $D; mkdir -p $D
tar --exclude=./.git --exclude=./gpurun_out --exclude='./_v*' --exclude=./profiles --exclude='*.o' -cf - . | tar -xf - -C $D
for f in $(git ls-tree --name-only $R paper_conf_icde_wei0l0lzj024_b200/csrc/); do git show $R:$f > $D/$f; done
(cd $D && python -c "
import importlib.util
spec = importlib.util.spec_from_file_location('b', 'paper_conf_icde_wei0l0lzj024_b200/build.py')
b = importlib.util.module_from_spec(spec); spec.loader.exec_module(b)
b.build(force=True)
")
echo "$D built from $R csrc/"
