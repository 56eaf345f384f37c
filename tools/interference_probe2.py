import torch
side = torch.cuda.Stream()
NB = 1 << 30
host_pin = torch.empty(NB, dtype=torch.uint8).pin_memory()
dev_big = torch.empty(NB, dtype=torch.uint8, device='cuda')
def ev_time(fn, reps=9):
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        fn(a, b)
        b.synchronize()
        out.append(a.elapsed_time(b) * 1e3)
    out.sort(); return round(out[len(out)//2], 1)
small = torch.zeros(1024, device='cuda')
for mib in (0, 24.5, 98, 392):
    n = max(int(mib * (1 << 18)), 1024)
    x = torch.ones(n, dtype=torch.int32, device='cuda'); y = torch.empty_like(x)
    def k(): torch.add(x, 1, out=y)
    def alone(a, b):
        torch.cuda._sleep(20000); a.record(); k(); b.record()
    def with_copy(d):
        def f(a, b):
            with torch.cuda.stream(side):
                if d == 'd2h': host_pin.copy_(dev_big, non_blocking=True)
                else: dev_big.copy_(host_pin, non_blocking=True)
            torch.cuda._sleep(20000); a.record(); k(); b.record()
            torch.cuda.synchronize()
        return f
    def many(d):
        # 10 back-to-back kernels during the copy
        def f(a, b):
            with torch.cuda.stream(side):
                host_pin.copy_(dev_big, non_blocking=True) if d == 'd2h' else dev_big.copy_(host_pin, non_blocking=True)
            torch.cuda._sleep(20000); a.record()
            for _ in range(10): k()
            b.record(); torch.cuda.synchronize()
        return f
    def many_alone(a, b):
        torch.cuda._sleep(20000); a.record()
        for _ in range(10): k()
        b.record()
    print(mib, 'add kernel us: alone', ev_time(alone), 'd2h', ev_time(with_copy('d2h')), 'h2d', ev_time(with_copy('h2d')),
          '| x10 alone', ev_time(many_alone), 'd2h', ev_time(many('d2h')), 'h2d', ev_time(many('h2d')))
