#!/bin/bash
# build locally (abort on failure), then run the given command on the B200 via gpurun
set -e
cd /root/repo
python -c "from paper_conf_sc_cui0czlzsmylg21_b200 import _build; _build.build()"
TIMEOUT=${GPU_TIMEOUT:-1500}
exec /usr/local/graft/bin/gpurun --timeout $TIMEOUT -- "$@"
