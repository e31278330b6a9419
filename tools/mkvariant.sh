#!/bin/bash
# tools/mkvariant.sh NAME "NVCC FLAGS..."  -> _vNAME/: a copy of the repo's python + sources with
# libltpg.so built with the extra flags (e.g. "-DLTPG_EXEC_MINB=5"); ships with gpurun for A/Bs
# (tools/ab.sh _vA _vB WORKLOAD...).
set -e
N=$1; F=$2
D=_v$N
rm -rf $D; mkdir -p $D
tar --exclude=./.git --exclude=./gpurun_out --exclude='./_v*' --exclude=./profiles --exclude='*.o' -cf - . | tar -xf - -C $D
(cd $D && python -c "
import importlib.util, sys
spec = importlib.util.spec_from_file_location('b', 'paper_conf_icde_wei0l0lzj024_b200/build.py')
b = importlib.util.module_from_spec(spec); spec.loader.exec_module(b)
b.build(force=True, extra=sys.argv[1].split())
" "$F")
echo "$D built with: $F"
