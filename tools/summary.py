import json,sys
for f in sys.argv[1:]:
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, 'ERR', e); continue
    print('==', f, 'value %.1f ms/step %.4f launches %s' % (d['value'], d['ms_per_step'], d['gpu_launches']))
    r=d['reroot']; print('  reroot sets', r['sets'], r['sets_original'], 'step_speedup', r['step_speedup'], 'UP speedup', r['updatePartials_speedup'])
    u=d['updatePartials']; print('  UP ms %.4f gflops %.1f share %.2f' % (u['ms_per_pass'], u['gflops'], u['share_of_step']))
    f_=d['roofline']; print('  roof achieved %.1f frac %.3f' % (f_['achieved'], f_['frac']))
    print('  e2e %.1f' % d['e2e']['value'], 'clk', d['clocks'])
