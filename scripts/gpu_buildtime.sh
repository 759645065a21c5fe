python -c "import __graft_entry__ as g; g.build()"
TM_TRACE_BUILD=1 timeout 2000 python -c "
import sys, time; sys.path.insert(0,'.')
import tmgen, paper_conf_eurosys_rogorapkmcc17_b200 as tmb
t=time.time(); wl=tmgen.config('${1:-C3}'); print('gen', round(time.time()-t,1), flush=True)
for ro in (0, 1):
    t=time.time(); db=tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=200000, tile_filter=1, row_order=ro); st=db.stats(); print('build row_order', ro, round(time.time()-t,2), 's', st['n_partitions'], 'partitions', st['n_rows'], 'rows', flush=True); db.close()
" 2>&1 | grep -v "^\[tm_build\] encode"
TM_FULL_SIZE=${1:-C3} timeout 3000 python -m pytest tests/test_gpu_full.py -m gpu -x -q -s 2>&1 | tail -9
