# usage: bash tools/gpu_ab.sh CFG ENGINE LIB... (runs tools/ab.py on the GPU box)
cd $GRAFT_REPO_ROOT
cfg=$1; eng=$2; shift 2
timeout 1500 python tools/ab.py $cfg $eng "$@" 2>&1 | tail -n $(( $# + 2 ))
