# variants on C2 (correctness subset + bench) then an ncu capture of the first one
# usage: bash scripts/gpu_var_prof.sh <tag> "<variants>"
TAG=$1; VARS=${2:-"5 0 2"}
bash scripts/gpu_variants.sh "$VARS" C2
bash scripts/gpu_profile_var.sh $TAG ${VARS%% *}
