# build libtg.so with extra nvcc flags for one source and keep it as variants/libtg_<name>.so
# (select at run time with TG_LIB=variants/libtg_<name>.so); rebuild the default afterwards
name=$1; src=$2; shift 2
env TG_EXTRA_FLAGS_${src^^}="$*" python -c "from paper_conf_ppopp_wangm23_b200.build import build; build(force=True)" || exit 1
mkdir -p variants; cp paper_conf_ppopp_wangm23_b200/libtg.so variants/libtg_$name.so
